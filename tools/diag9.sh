cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for t in 0 1; do echo "== BDL_GEN_TMA=$t"; for c in cfg4 cfg3; do BDL_GEN_TMA=$t timeout 200 python tools/time_subgraphs.py $c; done; done
timeout 200 python tools/gen_prof.py cfg4 4 7 26
