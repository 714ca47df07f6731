# per-kernel device times of one reduce step (ncu, serialised) + the bench line
NCU=/usr/local/cuda/bin/ncu
$NCU --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches.csv python tools/prof_step.py --warmup 1 --steps 1 > /dev/null 2>&1
python - <<'PY'
import csv
rows=list(csv.reader(open('gpurun_out/launches.csv')))
hdr=next(i for i,r in enumerate(rows) if 'Kernel Name' in r); h=rows[hdr]
ki,vi=h.index('Kernel Name'),h.index('Metric Value')
lst=[(r[ki].split('(')[0].split('::')[-1], float(r[vi])/1e3) for r in rows[hdr+1:] if len(r)>vi]
n=len(lst)//2 if len(lst)>4 else len(lst)
step=[x for x in lst[2:]][len(lst[2:])//2:]
print(' '.join(f'{k}={v:.1f}us' for k,v in step), '| total', round(sum(v for _,v in step),1))
PY
python bench.py --steps 5 --warmup 3 --no-cpu-baseline 2>&1 | tail -1 | python -c "import json,sys;d=json.loads(sys.stdin.read());print('bench', round(d['value']/1e9,2), 'G rec/s', round(d['ms_per_step'],3), 'ms')"
