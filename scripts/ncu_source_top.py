import csv, sys, subprocess
f=sys.argv[1]; n=int(sys.argv[2]) if len(sys.argv)>2 else 40
out=subprocess.run(['ncu','-i',f,'--page','source','--csv','--print-source','sass'],capture_output=True,text=True).stdout
rows=list(csv.reader(out.splitlines()))
hdr=rows[1]; data=rows[2:]
iS=hdr.index('Warp Stall Sampling (All Samples)'); iI=hdr.index('Instructions Executed'); iSrc=hdr.index('Source'); iA=hdr.index('Address')
tot=sum(int(r[iS]) for r in data if r[iS].isdigit()); toti=sum(int(r[iI]) for r in data if r[iI].isdigit())
print('samples',tot,'inst',toti,'ninstr',len(data))
mode=sys.argv[3] if len(sys.argv)>3 else 'stall'
key=(lambda r:-int(r[iS]) if r[iS].isdigit() else 0) if mode=='stall' else (lambda r:-int(r[iI]) if r[iI].isdigit() else 0)
for i,r in enumerate(data):
    r.append(i)
top=sorted(data,key=key)[:n]
for r in sorted(top,key=lambda r:r[-1]): print(r[-1], r[iS], r[iI], r[iSrc][:90])
