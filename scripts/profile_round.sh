#!/bin/bash
# Run on the GPU box (gpurun): launch list of the bench command + ncu --set full of the CPU-Free
# kernels (20/21-iteration launches) for C2 (time-blocked K=5 default, K=2), C2 per-iteration, C3 per-iteration and
# C3 time-blocked (K=3), under gpurun_out/.
set -x
out=gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches_c2.csv \
    python bench.py --steps 2 --warmup 3 > $out/launches_c2.log 2>&1
run_full() {  # name, kernel regex, bench args
  ncu --set full --clock-control none --import-source on -k "regex:$2" -c 1 \
      -o $out/full_$1 python bench.py --no-extras --steps 1 --warmup 3 --iters 20 ${@:3} > $out/full_$1.log 2>&1
  ncu -i $out/full_$1.ncu-rep --page raw --csv > $out/full_$1_raw.csv 2>/dev/null
  ncu -i $out/full_$1.ncu-rep --page details --csv > $out/full_$1_details.csv 2>/dev/null
}
run_full c2_tblock jb_tblock --config c2
run_full c2_tblock_k2 jb_tblock --config c2 --param tb_k=2
run_full c2 jb_sweep --config c2 --param tblock=0
run_full c3 jb_sweep --config c3 --param tblock=0
run_full c3_tblock jb_tblock --config c3 --iters 21
