#!/bin/bash
# End-of-round evidence on one B200 (under gpurun): smoke, the GPU suite, tools/round_evidence.sh
# (bench lines + launch lists), and one `ncu --set full` capture of a C5 bulk update launch.
mkdir -p gpurun_out/ev
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/ev/smoke.log 2>&1; echo "smoke rc=$?" >> gpurun_out/ev/smoke.log
timeout 1500 python -m pytest tests -m gpu -q > gpurun_out/ev/gpu_tests.log 2>&1; echo "tests rc=$?" >> gpurun_out/ev/gpu_tests.log
bash tools/round_evidence.sh
B="python bench.py --steps 1 --warmup 1 --no-e2e --no-cpu-baseline"
$B > gpurun_out/ev/plain_C5.log 2>&1 && \
timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled \
    -k "regex:update_kernel16<.int.512, .int.32>" -s 8 -c 1 -o /tmp/upd_C5 $B > gpurun_out/ev/ncu_full_C5.log 2>&1 && \
ncu -i /tmp/upd_C5.ncu-rep --page raw --csv > gpurun_out/ev/upd_C5_raw.csv && \
ncu -i /tmp/upd_C5.ncu-rep --page source --csv --print-source sass > gpurun_out/ev/upd_C5_src.csv
tail -2 gpurun_out/ev/gpu_tests.log; tail -1 gpurun_out/ev/smoke.log
