#!/bin/bash
# Run on the GPU box (gpurun): bench line + launch list + one ncu --set full
# capture of the dominant kernel for one workload.  Usage:
#   scripts/profile.sh <tag> <algo> <config> [extra bench args]
set -u
tag=$1; algo=$2; cfg=$3; shift 3
out=gpurun_out
mkdir -p $out
timeout 900 python bench.py --algo $algo --config $cfg "$@" > $out/${tag}_bench.json 2> $out/${tag}_bench.log
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/${tag}_launches.csv \
    python bench.py --algo $algo --config $cfg --no-extras --steps 2 --warmup 3 "$@" > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:path_kernel -s 3 -c 1 \
    -o $out/${tag} python bench.py --algo $algo --config $cfg --no-extras --steps 1 --warmup 3 "$@" > $out/${tag}_ncu.log 2>&1
tail -2 $out/${tag}_ncu.log
