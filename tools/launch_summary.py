import csv, collections, sys
rows=list(csv.reader(open(sys.argv[1])))
hi=[i for i,r in enumerate(rows) if 'Kernel Name' in r][0]
h=rows[hi]; ki=h.index('Kernel Name'); vi=h.index('Metric Value')
data=[(r[ki], float(r[vi].replace(',',''))) for r in rows[hi+1:] if len(r)>vi]
# keep only the last step's worth: identify by k_adam occurrences
names=[k.split('(')[0].split('<')[0].replace('void ','') for k,_ in data]
idx=[i for i,n in enumerate(names) if n.endswith('k_adam')]
lo = idx[-2]+1 if len(idx)>=2 else 0; hi2 = idx[-1]+1
agg=collections.defaultdict(lambda:[0,0.0])
for n,(k,v) in zip(names[lo:hi2], data[lo:hi2]):
    agg[n][0]+=1; agg[n][1]+=v
tot=sum(v for _,v in agg.values())
print(f"one step (launches {lo}..{hi2-1}): {hi2-lo} launches, {tot/1e6:.3f} ms serialised")
for k,(n,v) in sorted(agg.items(), key=lambda x:-x[1][1]): print(f"{k:32s} {n:4d} {v/1e3:9.1f} us {100*v/tot:5.1f}%")
