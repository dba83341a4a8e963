import csv,collections,sys,subprocess,io
rep=sys.argv[1]
txt=subprocess.run(['ncu','-i',rep,'--page','details','--csv'],capture_output=True,text=True).stdout
r=list(csv.reader(io.StringIO(txt))); h=r[0]
for x in r[1:]:
    n=x[h.index('Metric Name')]
    if n in ['Duration','Executed Instructions','Issue Slots Busy','Registers Per Thread','Achieved Active Warps Per SM','Eligible Warps Per Scheduler','DRAM Throughput','L1/TEX Hit Rate','Mem Busy','Max Bandwidth']:
        print(n, x[h.index('Metric Value')], x[h.index('Metric Unit')])
txt=subprocess.run(['ncu','-i',rep,'--page','source','--csv','--print-source','sass'],capture_output=True,text=True).stdout
rows=list(csv.reader(io.StringIO(txt)))
hdr=rows[1]; ix={h:i for i,h in enumerate(hdr)}
data=[r for r in rows[2:] if len(r)==len(hdr)]
ie=ix['Instructions Executed']
ops=collections.Counter(); n=0
for r in data:
    v=int(r[ie] or 0); n+=v
    s=r[ix['Source']].split(); op=s[1] if s[0].startswith('@') else s[0]
    ops[op.split('.')[0]]+=v
print(n, ' '.join(f'{k}:{v/1e6:.2f}' for k,v in ops.most_common(22)))
scols=[h for h in hdr if h.startswith('stall_') and 'Not Issued' not in h]
tot=collections.Counter()
for r in data:
    for h in scols: tot[h]+=float(r[ix[h]] or 0)
s=sum(tot.values())
print([(k[6:],round(100*v/s,1)) for k,v in tot.most_common(10)])
