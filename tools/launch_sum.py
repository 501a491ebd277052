"""Sum an ncu --csv launch list (gpu__time_duration.sum) by kernel: python tools/launch_sum.py list.csv [top]"""
import collections
import csv
import io
import sys

U = {'nsecond': 1e-3, 'usecond': 1, 'msecond': 1e3, 'ns': 1e-3, 'us': 1, 'ms': 1e3}
txt = open(sys.argv[1]).read()
rows = list(csv.DictReader(io.StringIO(txt[txt.index('"ID"'):])))
agg = collections.OrderedDict()
for r in rows:
    if r['Metric Name'] != 'gpu__time_duration.sum':
        continue
    k = r['Kernel Name'][:90]
    v = float(r['Metric Value'].replace(',', '')) * U[r['Metric Unit']]
    agg.setdefault(k, [0, 0])
    agg[k][0] += v
    agg[k][1] += 1
print('total us', round(sum(v[0] for v in agg.values())))
for k, v in sorted(agg.items(), key=lambda x: -x[1][0])[:int(sys.argv[2]) if len(sys.argv) > 2 else 12]:
    print('  %8.0f %4d %s' % (v[0], v[1], k))
