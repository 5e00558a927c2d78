cd $GRAFT_REPO_ROOT
timeout 300 python -m pytest tests/test_gpu_gen.py tests/test_gpu_parity.py -x -q 2>&1 | tail -2
for c in cfg5 cfg4 cfg3; do for r in _ab/head . _ab/head .; do timeout 120 python tools/ab_sub.py $r $c; done; done
