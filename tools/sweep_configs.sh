cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
for c in cfg1 cfg2 cfg5 cfg3 cfg4; do
  timeout 400 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/sweep_$c.json 2> gpurun_out/sweep_$c.err
  echo "$c rc=$?"; tail -c 600 gpurun_out/sweep_$c.json
done
