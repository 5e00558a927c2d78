cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests/test_gpu_sharding.py -x -q 2>&1 | tail -5
timeout 300 python bench.py --config cfg5 --spatial --steps 5 --warmup 3 2>&1 | tail -2
