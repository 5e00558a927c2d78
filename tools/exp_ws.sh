for cfg in "BDL_LAG=9" "BDL_LAG=9 BDL_WS_DBG=1" "BDL_LAG=9 BDL_WS_DBG=2" "BDL_LAG=9 BDL_WS_DBG=3"; do
  echo "== $cfg"; env $cfg python tools/trace_ws.py memoized 2>&1 | grep -E "kernel ms|load |mma |epilogue|cta_span"
done
