#!/bin/bash
# Final round-2 validation on the GPU box (gpurun): GPU test suite, smoke, bench lines of every
# config (+ virtual-slab lines, the reference arm), the C5 latency sweep, and the launch list of
# the default bench command — all under gpurun_out/ (prefix f_; re-run as the last validation of the round).
out=gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.limit,temperature.gpu --format=csv > $out/f_smi.txt
timeout 1200 python -m pytest tests -m gpu -q > $out/f_pytest_gpu.log 2>&1; echo "rc=$?" >> $out/f_pytest_gpu.log
python -c "import __graft_entry__ as g; g.smoke()" > $out/f_smoke.log 2>&1; echo "rc=$?" >> $out/f_smoke.log
python bench.py > $out/f_bench_c2.json 2> $out/f_bench_c2.err
for c in c1 c3 c4 c5a c5b; do python bench.py --config $c > $out/f_bench_$c.json 2> $out/f_bench_$c.err; done
python bench.py --no-extras --virtual 8 > $out/f_bench_c2_v8.json 2> $out/f_bench_c2_v8.err
python bench.py --no-extras --config c3 --virtual 2 > $out/f_bench_c3_v2.json 2> $out/f_bench_c3_v2.err
python bench.py --impl reference > $out/f_bench_reference.json 2> $out/f_bench_reference.err
timeout 1200 python bench_latency.py --out $out/f_latency_sweep.json > $out/f_latency.log 2>&1
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/f_launches_c2.csv \
    python bench.py --steps 2 --warmup 3 > $out/f_launches_c2.log 2>&1
