cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
timeout 300 python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err; echo bench rc=$?; tail -c 3000 gpurun_out/bench_default.json
for c in cfg1 cfg5 cfg3 cfg4; do
  timeout 400 python bench.py --config $c --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/sweep_$c.json 2> gpurun_out/sweep_$c.err
  echo "$c rc=$?"; tail -c 1500 gpurun_out/sweep_$c.json
done
