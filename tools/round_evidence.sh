#!/bin/bash
# Round evidence on one B200 (run under gpurun): bench lines for every config, the FP32 C5 line,
# the least-squares line, the reference (oracle) arm, a 2-rank multi-process bench (ranks share the
# GPU: a plumbing check), and the ncu launch lists of the bench command (C5, C4).  -> gpurun_out/ev/
mkdir -p gpurun_out/ev
for c in C1 C2 C3 C4; do
  timeout 600 python bench.py --config $c > gpurun_out/ev/bench_$c.json 2> gpurun_out/ev/bench_$c.err
done
timeout 900 python bench.py > gpurun_out/ev/bench_C5.json 2> gpurun_out/ev/bench_C5.err
timeout 900 python bench.py --dtype f32 > gpurun_out/ev/bench_C5_f32.json 2> gpurun_out/ev/bench_C5_f32.err
timeout 900 python bench.py --solve 4736 --no-e2e --no-cpu-baseline > gpurun_out/ev/bench_C5_solve.json 2>&1
timeout 900 python bench.py --impl reference > gpurun_out/ev/bench_ref_C5.json 2>&1
timeout 900 python bench.py --gpus 2 --config C3 --no-cpu-baseline > gpurun_out/ev/bench_C3_g2.json 2> gpurun_out/ev/bench_C3_g2.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev/launches_C5.csv \
    python bench.py --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ev/ncu_launch_C5.log 2>&1
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ev/launches_C4.csv \
    python bench.py --config C4 --steps 1 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ev/ncu_launch_C4.log 2>&1
for f in gpurun_out/ev/bench_*.json; do echo "$f: $(tail -c 300 $f)"; done
