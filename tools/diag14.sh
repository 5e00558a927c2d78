cd $GRAFT_REPO_ROOT
for r in _ab/bf73d49 _ab/f654848 . _ab/bf73d49 .; do timeout 60 python tools/ab_ws.py $r; done
