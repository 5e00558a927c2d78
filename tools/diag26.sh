cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q 2>&1 | tail -3
timeout 120 python tools/ab_sub.py . cfg5
timeout 900 python tools/sweep_fig10_11.py 2>&1 | tee gpurun_out/r01c_fig10_11.txt
