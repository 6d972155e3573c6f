for v in final batch final batch; do JACOBI_LIB=$PWD/scratch/ab/$v.so timeout 300 python scripts/scope_ab.py --slabs 2,4 --out gpurun_out/v36_$v.jsonl > /dev/null 2>&1; python -c "
import json
for l in open('gpurun_out/v36_$v.jsonl'):
    r=json.loads(l)
    if r['no_compute'] and r['variant']!='cpufree_sys': print('$v', r['config'][:3], r['P'], r['variant'], r['us_per_iter'])
" >> gpurun_out/v36_summary.txt; done
JACOBI_LIB=$PWD/scratch/ab/batch.so timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_ll.py -m gpu -q > gpurun_out/v36_pytest.log 2>&1; echo rc=$? >> gpurun_out/v36_pytest.log
