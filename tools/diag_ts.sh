cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
BDL_TS=1 timeout 200 python tools/ws_dbg_sweep.py 0 2 8 2>&1 | grep median
BDL_TS=1 timeout 100 python tools/ts_prof.py 2>&1 | tail -8
BDL_TS=1 timeout 300 python -m pytest tests/test_gpu_parity.py -x -q 2>&1 | tail -3
