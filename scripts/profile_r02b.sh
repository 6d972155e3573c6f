#!/bin/bash
# Final ncu --set full capture of the C2 time-blocked kernel (hoisted shuffles), 20 iterations,
# raw / details / source pages under gpurun_out/ (prefix r02b_).
out=gpurun_out
ncu --set full --clock-control none --import-source on -k "regex:jb_tblock" -c 1 \
    -o $out/r02b_full_c2_tblock python bench.py --no-extras --steps 1 --warmup 3 --iters 20 --config c2 > $out/r02b_full_c2_tblock.log 2>&1
ncu -i $out/r02b_full_c2_tblock.ncu-rep --page raw --csv > $out/r02b_full_c2_tblock_raw.csv 2>/dev/null
ncu -i $out/r02b_full_c2_tblock.ncu-rep --page details --csv > $out/r02b_full_c2_tblock_details.csv 2>/dev/null
ncu -i $out/r02b_full_c2_tblock.ncu-rep --page source --csv > $out/r02b_full_c2_tblock_source.csv 2>/dev/null
rm -f $out/r02b_full_c2_tblock.ncu-rep
