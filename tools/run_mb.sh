cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -std=c++17 -o /tmp/mma_mb tools/mma_microbench.cu && timeout 120 /tmp/mma_mb
timeout 600 python -m pytest tests -m gpu -x -q -k "gen or pool or parity" 2>&1 | tail -3
for c in cfg3 cfg4; do timeout 300 python bench.py --config $c --steps 3 --warmup 3 --no-cpu-baseline --no-cudnn 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$c', d['value'], d['ms_per_step'], d['roofline']['frac'])"; done
