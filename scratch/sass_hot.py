import csv, sys
r=list(csv.reader(open(sys.argv[1])))
n=int(sys.argv[2]) if len(sys.argv)>2 else 45
# first kernel section only
sec=[]; started=False
for row in r:
    if row and row[0]=='Kernel Name':
        if started: break
        started=True; continue
    sec.append(row)
h=sec[0]; body=sec[1:]
i=h.index('Warp Stall Sampling (All Samples)'); s=h.index('Source'); e=h.index('Instructions Executed')
f=lambda v: float(v) if v not in ('','-') else 0.0
tot=sum(f(x[i]) for x in body); toti=sum(f(x[e]) for x in body)
print("total inst", toti, "samples", tot, len(body))
rows=sorted(enumerate(body), key=lambda x:-f(x[1][e]))[:n]
for k,x in sorted(rows):
    print(k, x[e], x[i], x[s][:90])
