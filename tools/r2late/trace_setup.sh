cd $GRAFT_REPO_ROOT; O=gpurun_out/r2late; mkdir -p $O
AMGT_TRACE=1 python tools/r2late/setup_time.py cfg3 1 > $O/trace_setup.log 2>&1
python - <<'PY'
import re
enq=dev=0; rows=[]
for l in open('gpurun_out/r2late/trace_setup.log'):
    m=re.match(r'trace (.{20}) enqueue\s+(-?[\d.]+) ms\s+device-done\s+([\d.]+) ms', l)
    if m: rows.append((m.group(1).strip(), float(m.group(2)), float(m.group(3))))
n=len(rows)//2
last=rows[n:] if len(rows)%2==0 else rows
import collections
agg=collections.defaultdict(lambda:[0,0.0,0.0])
for name,e,d in last:
    a=agg[name]; a[0]+=1; a[1]+=max(e,0); a[2]+=d
tot_e=sum(a[1] for a in agg.values()); tot_d=sum(a[2] for a in agg.values())
print(f"segments {len(last)} host enqueue {tot_e:.2f} ms device {tot_d:.2f} ms")
for k,a in sorted(agg.items(), key=lambda x:-x[1][1])[:14]: print(f"  {k:20s} n={a[0]:3d} enqueue {a[1]:7.3f} ms device {a[2]:7.3f} ms")
PY
