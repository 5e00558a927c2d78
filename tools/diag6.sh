cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for c in cfg5 cfg4 cfg3; do timeout 200 python tools/time_subgraphs.py $c; done
