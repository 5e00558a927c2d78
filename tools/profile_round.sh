#!/bin/bash
# Round profiling: launch list (cold, serialized) + one full ncu capture of each hot kernel.
# Usage (under gpurun): bash tools/profile_round.sh r01
R=${1:-r01}
mkdir -p gpurun_out
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 60 --csv \
    --log-file gpurun_out/${R}_launches.csv python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-cudnn > /dev/null 2>&1
echo launches=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:memo_ws -s 3 -c 1 \
    -o gpurun_out/${R}_memo_ws python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-cudnn > /dev/null 2>&1
echo memo=$?
timeout 600 ncu --set full --clock-control none -k regex:brickify -s 2 -c 2 \
    -o gpurun_out/${R}_brickify python bench.py --steps 1 --warmup 3 --no-cpu-baseline --no-cudnn > /dev/null 2>&1
echo brickify=$?
timeout 600 ncu --set full --clock-control none -k regex:tc_padded -s 1 -c 1 \
    -o gpurun_out/${R}_padded python bench.py --steps 1 --warmup 3 --mode padded --no-cpu-baseline --no-cudnn > /dev/null 2>&1
echo padded=$?
timeout 600 ncu --set full --clock-control none --import-source on -k regex:gen_kernel -s 1 -c 1 \
    -o gpurun_out/${R}_gen_cfg5 python bench.py --config cfg5 --steps 1 --warmup 3 --no-cpu-baseline --no-cudnn > /dev/null 2>&1
echo gen_cfg5=$?
for c in cfg3 cfg4; do
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none -c 200 --csv \
      --log-file gpurun_out/${R}_launches_$c.csv python bench.py --config $c --steps 1 --warmup 3 --no-cpu-baseline --no-cudnn > /dev/null 2>&1
  echo launches_$c=$?
done
