cd $GRAFT_REPO_ROOT
timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for c in cfg4 cfg3; do for r in _ab/head . _ab/head .; do timeout 120 python tools/ab_sub.py $r $c; done; done
timeout 200 python tools/time_subgraphs.py cfg4 | grep -E "padded|total"
timeout 200 python tools/time_subgraphs.py cfg3 | grep -E "padded|total"
