#!/bin/bash
# Run on the GPU box: bench line, ncu launch list of the bench command, ncu --set full of the
# dominant (bulk update) kernel.  Outputs land in gpurun_out/ (copy summaries to profiles/).
set -x
CFG=${CFG:-C5}
timeout 600 python bench.py --config $CFG > gpurun_out/bench_$CFG.json 2> gpurun_out/bench_$CFG.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$CFG.csv \
    python bench.py --config $CFG --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_launch_$CFG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:update_kernel -s 1 -c 1 \
    -o gpurun_out/full_update_$CFG python bench.py --config $CFG --steps 1 --warmup 3 --no-e2e --no-cpu-baseline \
    > gpurun_out/ncu_full_$CFG.log 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:panel_kernel -s 1 -c 1 \
    -o gpurun_out/full_panel_$CFG python bench.py --config $CFG --steps 1 --warmup 3 --no-e2e --no-cpu-baseline \
    > gpurun_out/ncu_fullp_$CFG.log 2>&1
ls -la gpurun_out
