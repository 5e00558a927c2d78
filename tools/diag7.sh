cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for rep in 1 2; do for d in 0 1 2 3; do echo "== dbg $d"; BDL_GEN_DBG=$d timeout 200 python tools/time_subgraphs.py cfg4 | grep -E "total|\[14,14\]|\[46,46\]"; BDL_GEN_DBG=$d timeout 200 python tools/time_subgraphs.py cfg5 | grep total; done; done
