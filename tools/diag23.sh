cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for c in cfg5 cfg3 cfg4; do BDL_GEN_GEOM=1 timeout 120 python tools/time_subgraphs.py $c --reps 3 2>&1 | grep -v "^gen sg" ; done
BDL_GEN_GEOM=1 timeout 120 python tools/time_subgraphs.py cfg5 --reps 1 2>&1 | grep "gen sg" | head -2
for c in cfg5 cfg3 cfg4; do for r in _ab/head . ; do timeout 120 python tools/ab_sub.py $r $c; done; done
