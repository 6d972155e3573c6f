#!/bin/bash
# Run on the GPU box (gpurun): launch list of the bench command + ncu --set full of the
# persistent kernel for C2 and C3 (20-iteration launches), outputs under gpurun_out/.
set -x
out=gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches_c2.csv \
    python bench.py --steps 2 --warmup 3 > $out/launches_c2.log 2>&1
for cfg in c2 c3; do
  ncu --set full --clock-control none --import-source on -k regex:jb_sweep -c 1 \
      -o $out/full_$cfg python bench.py --config $cfg --no-extras --steps 1 --warmup 3 --iters 20 \
      > $out/full_$cfg.log 2>&1
  ncu -i $out/full_$cfg.ncu-rep --page raw --csv > $out/full_${cfg}_raw.csv 2>/dev/null
  ncu -i $out/full_$cfg.ncu-rep --page details --csv > $out/full_${cfg}_details.csv 2>/dev/null
done
