import csv, sys, subprocess
f=sys.argv[1]; step=int(sys.argv[2]) if len(sys.argv)>2 else 50
out=subprocess.run(['ncu','-i',f,'--page','source','--csv','--print-source','sass'],capture_output=True,text=True).stdout
rows=list(csv.reader(out.splitlines()))
hdr=rows[1]; data=rows[2:]
iS=hdr.index('Warp Stall Sampling (All Samples)'); iI=hdr.index('Instructions Executed'); iSrc=hdr.index('Source')
for b in range(0,len(data),step):
    seg=data[b:b+step]
    ins=sum(int(r[iI]) for r in seg if r[iI].isdigit()); st=sum(int(r[iS]) for r in seg if r[iS].isdigit())
    if ins>0.01*sum(int(r[iI]) for r in data if r[iI].isdigit()) or st>50:
        first=[r[iSrc].strip()[:40] for r in seg[:3]]
        print(b, ins, st, first)
