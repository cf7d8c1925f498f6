for i in 1 2 3; do echo "W16"; TQR_W16=1 bash tools/quickbench.sh C5 C3; echo "BASE"; bash tools/quickbench.sh C5 C3; done > gpurun_out/exp_ab.txt 2>&1
cat gpurun_out/exp_ab.txt
