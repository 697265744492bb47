import csv, sys
rows=list(csv.DictReader(l for l in open(sys.argv[1]) if not l.startswith('==')))
idx=[i for i,r in enumerate(rows) if 'set_step_kernel' in r['Kernel Name']]
k=int(sys.argv[2]) if len(sys.argv)>2 else len(idx)//2
a,b=idx[k],idx[k+1]
tot=0
for r in rows[a:b]:
    v=float(r['Metric Value'].replace(',',''));u=r['Metric Unit']
    v*={'nsecond':1,'ns':1,'usecond':1e3,'us':1e3,'msecond':1e6}.get(u,1)
    tot+=v
    print(f"{v/1e3:8.1f} {r['Kernel Name'][:70]}")
print(f"{tot/1e3:.1f} us serialised")
