cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 200 python tools/time_subgraphs.py cfg4
timeout 200 python tools/time_subgraphs.py cfg4 --mode memoized
