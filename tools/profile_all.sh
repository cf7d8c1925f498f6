#!/bin/bash
# Round-end evidence run on the GPU box (outputs in gpurun_out/, summaries copied to profiles/).
set -x
python -c "import __graft_entry__ as g; g.build(); g.smoke()" > gpurun_out/smoke.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_C5.json 2> gpurun_out/bench_C5.err
timeout 900 python bench.py --dtype f32 > gpurun_out/bench_C5_f32.json 2> gpurun_out/bench_C5_f32.err
for c in C1 C2 C3 C4; do timeout 600 python bench.py --config $c --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err; done
timeout 600 python bench.py --impl reference --steps 1 --warmup 0 > gpurun_out/bench_ref_C5.json 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_C5.csv \
    python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_C5_f32.csv \
    python bench.py --dtype f32 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:update_kernel -s 8 -c 1 \
    -o gpurun_out/full_update_C5 python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:update_kernel32 -s 8 -c 1 \
    -o gpurun_out/full_update32_C5 python bench.py --dtype f32 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:domain_kernel -s 2 -c 1 \
    -o gpurun_out/full_domain_C4 python bench.py --config C4 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1
ls -la gpurun_out
