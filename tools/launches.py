import csv, collections, sys
f=sys.argv[1]; steps=int(sys.argv[2]) if len(sys.argv)>2 else 1
rows=list(csv.DictReader(l for l in open(f) if not l.startswith('==')))
agg=collections.defaultdict(lambda:[0,0.0])
for r in rows:
    n=r['Kernel Name'][:80]; v=float(r['Metric Value'].replace(',',''))
    u=r['Metric Unit']; v*= {'nsecond':1,'ns':1,'usecond':1e3,'us':1e3,'msecond':1e6,'ms':1e6}.get(u,1)
    agg[n][0]+=1; agg[n][1]+=v
tot=sum(v for _,v in agg.values())
print(f"total {tot/1e3:.1f} us over {len(rows)} launches")
for n,(c,v) in sorted(agg.items(), key=lambda x:-x[1][1])[:30]:
    print(f"{c:5d} {v/1e3/steps:9.1f}us/step {100*v/tot:5.1f}% {n}")
