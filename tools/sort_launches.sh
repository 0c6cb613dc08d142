ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv --log-file gpurun_out/sort_launches.csv python tools/bench_sort.py ${1:-13000000} > /dev/null 2>&1
python tools/bench_sort.py ${1:-13000000}
python - <<'PY'
import csv
from collections import defaultdict
lines=open("gpurun_out/sort_launches.csv").read().splitlines()
i=[k for k,l in enumerate(lines) if l.startswith('"ID"')][0]
rows=list(csv.reader(lines[i:])); h=rows[0]
d=defaultdict(dict); names={}
for r in rows[1:]:
    if len(r)<5: continue
    kid=int(r[h.index("ID")]); names[kid]=r[h.index("Kernel Name")][:30]; d[kid][r[h.index("Metric Name")]]=r[h.index("Metric Value")]
for kid in sorted(d)[-14:]:
    m=d[kid]; print(kid, names[kid], m.get('gpu__time_duration.sum'), 'rd',m.get('dram__bytes_read.sum'),'wr',m.get('dram__bytes_write.sum'))
PY
