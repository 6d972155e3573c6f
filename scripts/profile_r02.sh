#!/bin/bash
# Round-2 evidence on the GPU box (gpurun): launch list of the default bench command and
# ncu --set full captures of the CPU-Free kernels the benchmarks run (20/21-iteration launches):
# C2 time-blocked K = 5 (warp-specialised), C3 time-blocked K = 3 (warp-specialised), and the
# per-iteration streaming kernel for C2 — all under gpurun_out/.
set -x
out=gpurun_out
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/r02_launches_c2.csv \
    python bench.py --steps 2 --warmup 3 > $out/r02_launches_c2.log 2>&1
run_full() {  # name, kernel regex, bench args
  ncu --set full --clock-control none --import-source on -k "regex:$2" -c 1 \
      -o $out/r02_full_$1 python bench.py --no-extras --steps 1 --warmup 3 --iters 20 ${@:3} > $out/r02_full_$1.log 2>&1
  ncu -i $out/r02_full_$1.ncu-rep --page raw --csv > $out/r02_full_$1_raw.csv 2>/dev/null
  ncu -i $out/r02_full_$1.ncu-rep --page details --csv > $out/r02_full_$1_details.csv 2>/dev/null
  ncu -i $out/r02_full_$1.ncu-rep --page source --csv > $out/r02_full_$1_source.csv 2>/dev/null
}
run_full c2_tblock jb_tblock --config c2
run_full c3_tblock jb_tblock --config c3 --iters 21
run_full c2 jb_sweep --config c2 --param tblock=0
