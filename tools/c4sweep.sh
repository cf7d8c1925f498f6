python -m pytest tests/test_gpu_parity.py -q -x -k "tree or merge" > gpurun_out/pytest_tree.log 2>&1; tail -3 gpurun_out/pytest_tree.log
for g in -1 0 8 20 37; do bash tools/treesweep.sh C4 0 "--tree-group $g" | sed "s/^/G=$g /"; done
for sp in 1 4; do TQR_MERGE_SPLIT=$sp bash tools/treesweep.sh C4 0 | sed "s/^/split=$sp /"; done
