cd $GRAFT_REPO_ROOT
timeout 300 python -m pytest tests/test_gpu_gen.py tests/test_gpu_parity.py -x -q 2>&1 | tail -2
for c in cfg4 cfg3; do timeout 200 python tools/time_subgraphs.py $c | grep -E "cuda-core|\[ 0,|total"; done
