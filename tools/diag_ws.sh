cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python tools/ws_dbg_sweep.py 0 1 2 8 16 24 2>&1 | grep median
MODE=padded timeout 100 python tools/ws_dbg_sweep.py 0 2>&1 | grep median
timeout 120 python tools/trace_ws.py memoized 2>&1 | tail -14
