#!/bin/bash
# lookahead overlapped with its panel (default) vs after the panel (TQR_LA_OVERLAP=0)
timeout 900 python -m pytest tests -m gpu -q -x > gpurun_out/pytest_gpu.log 2>&1; tail -3 gpurun_out/pytest_gpu.log
for c in ${@:-C2 C3 C5}; do
  TQR_LA_OVERLAP=0 bash tools/quickbench.sh $c | sed 's/^/ovl=0 /'
  bash tools/quickbench.sh $c | sed 's/^/ovl=1 /'
done
