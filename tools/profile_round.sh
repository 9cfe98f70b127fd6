#!/bin/bash
# One GPU session: bench (tuned), then the ncu launch list of the bench command and --set full
# captures of the dominant hotspot kernel (bench granularity) and of srad_stream.  Outputs under
# gpurun_out/; tools/ncu_summary.py turns them into profiles/ summaries.
set -x
TAG=${1:-r01}
python bench.py > gpurun_out/bench_${TAG}.json 2> gpurun_out/bench_${TAG}.err
G=$(python -c "import json;print(','.join(map(str,json.load(open('gpurun_out/bench_${TAG}.json'))['config']['granularity'])))")
echo "tuned granularity: $G"
ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_${TAG}.csv \
    python bench.py --steps 1 --warmup 3 --gran $G --no-extra --no-cpu > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:hs_stream -s 12 -c 1 -o gpurun_out/prof_${TAG}_hotspot \
    python bench.py --steps 1 --warmup 3 --gran $G --no-extra --no-cpu --iters 48 > gpurun_out/ncu_${TAG}.log 2>&1
GS=$(python -c "import json;print(','.join(map(str,json.load(open('gpurun_out/bench_${TAG}.json'))['workloads']['srad']['tuned']['g'])))")
echo "srad tuned granularity: $GS"
ncu --set full --clock-control none --import-source on -k regex:srad_stream -s 3 -c 1 -o gpurun_out/prof_${TAG}_srad \
    python tools/prof_srad.py $GS > gpurun_out/ncu_${TAG}_srad.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}_srad.csv \
    python tools/prof_srad.py $GS > /dev/null 2>&1
tail -2 gpurun_out/ncu_${TAG}.log
# lud panel 128 (tensor-core trailing update): launch list of one factorisation + a full capture
# of the largest rank-128 update (the first one)
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_${TAG}_lud128.csv \
    python tools/prof_lud.py 8192 1,1,1,1,1,0,0 128 > /dev/null 2>&1
ncu --set full --clock-control none --import-source on -k regex:lud_tc -s 3 -c 1 -o gpurun_out/prof_${TAG}_lud128 \
    python tools/prof_lud.py 8192 1,1,1,1,1,0,0 128 > gpurun_out/ncu_${TAG}_lud128.log 2>&1
