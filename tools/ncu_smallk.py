import csv, collections, sys
rows=list(csv.reader(open(sys.argv[1])))
hi=next(i for i,r in enumerate(rows) if "Kernel Name" in r)
h=rows[hi]; ki=h.index("ID"); mi=h.index("Metric Name"); vi=h.index("Metric Value")
per=collections.OrderedDict()
for r in rows[hi+1:]:
    if len(r)>vi: per.setdefault(r[ki],{})[r[mi]]=r[vi]
vals=list(per.values())
for i, name in zip(range(20,len(vals),40), ("4K","64K","1M","4M","38.5M")):
    seg=vals[i:i+20]
    print(name, seg[0].get("launch__grid_size"), sorted(float(v["gpu__time_duration.sum"].replace(",","")) for v in seg)[len(seg)//2])
