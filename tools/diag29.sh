cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for v in 0 1 0 1; do BDL_GEN_SW64=$v timeout 120 python tools/ab_sub.py . cfg5; done
BDL_GEN_GEOM=1 timeout 120 python tools/time_subgraphs.py cfg5 --reps 1 2>&1 | grep "gen sg" | head -1
timeout 120 python tools/gen_prof.py cfg5
