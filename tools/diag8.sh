cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python -m pytest tests/test_gpu_gen.py -x -q 2>&1 | tail -2
timeout 200 python tools/gen_prof.py cfg5
timeout 200 python tools/gen_prof.py cfg4 0 2 3 4 6 7 13 14 26
timeout 200 python tools/gen_prof.py cfg3 0 1 4
