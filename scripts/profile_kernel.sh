#!/bin/bash
# One ncu --set full capture of a CPU-Free kernel launch under bench.py (GPU box, via gpurun):
#   scripts/profile_kernel.sh NAME KERNEL_REGEX [bench.py args]
# -> gpurun_out/NAME.ncu-rep and its raw / details / source pages as CSV.
out=gpurun_out
name=$1; rx=$2; shift 2
ncu --set full --clock-control none --import-source on -k "regex:$rx" -c 1 \
    -o $out/$name python bench.py --no-extras --steps 1 --warmup 3 "$@" > $out/$name.log 2>&1
ncu -i $out/$name.ncu-rep --page raw --csv > $out/${name}_raw.csv 2>/dev/null
ncu -i $out/$name.ncu-rep --page details --csv > $out/${name}_details.csv 2>/dev/null
ncu -i $out/$name.ncu-rep --page source --csv > $out/${name}_source.csv 2>/dev/null
