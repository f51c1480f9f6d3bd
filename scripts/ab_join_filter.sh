python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for v in 1 0 1 0; do LASAGNA_JOIN_FILTER=$v python bench.py --no-cpu-baseline --steps 5 > gpurun_out/ab_$v.log 2>&1; python -c "
import json; d=json.load(open('gpurun_out/ab_$v.log')); print('filter=$v', round(d['ms_per_step'],2), d['read_end_pairs'], {k:round(v['ms_per_step'],2) for k,v in d['roofline']['phases'].items()})" >> gpurun_out/ab.txt; done
