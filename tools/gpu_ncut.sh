ncu --metrics gpu__time_duration.sum,launch__grid_size,smsp__inst_executed.sum --clock-control none -k regex:"verify|compact|levels" -s 12 -c 8 --csv python tools/step_timeline.py > gpurun_out/ncut.csv 2>/dev/null
python3 - <<'PY'
import csv,collections
rows=list(csv.reader(open('gpurun_out/ncut.csv')))
hdr=None; d=collections.OrderedDict()
for r in rows:
    if r and r[0]=='ID': hdr=r; continue
    if hdr and len(r)==len(hdr):
        z=dict(zip(hdr,r)); d.setdefault((z['ID'],z['Kernel Name'][:40]),{})[z['Metric Name']]=z['Metric Value']
for k,v in d.items(): print(k, v)
PY
