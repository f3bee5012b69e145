import csv,sys
rows=list(csv.reader(open(sys.argv[1])))
hdr=None; out=[]
for r in rows:
    if r and r[0]=='ID': hdr=r; continue
    if hdr and len(r)==len(hdr):
        d=dict(zip(hdr,r))
        if d['Metric Name']=='gpu__time_duration.sum':
            v=float(d['Metric Value'].replace(',',''))
            if d['Metric Unit']=='ns': v/=1000
            out.append((d['Kernel Name'], d['Grid Size'], v))
tot=sum(x[2] for x in out)
for i,(k,g,t) in enumerate(out): print(i,k,g,round(t,2))
print("total us", round(tot,1))
