"""Instruction / stall split of a sampling kernel by code region, from an ncu source-page export
(`ncu -i rep --page source --csv --print-source cuda,sass > src.csv`).  Region line ranges refer to
gsword_kernels.cu at the profiled commit; device_util.cuh lines are listed separately.
usage: python scripts/ncu_regions.py "sample_kernel<(int)1" unused src.csv"""
import csv,collections,sys
rows=list(csv.reader(open(sys.argv[3] if len(sys.argv) > 3 else '/tmp/src_all.csv')))
kernel=None;hdr=None;data=collections.defaultdict(lambda: collections.defaultdict(lambda:[0,0,0,'']))
fileidx=0
for r in rows:
    if not r: continue
    if r[0]=="Function Name": kernel=r[1]; fileidx+=1; continue
    if r[0]=="Line No": hdr=r; continue
    if hdr and kernel and r[0].isdigit() and len(r)==len(hdr) and r[2]=="-":
        ie=hdr.index("Instructions Executed"); te=hdr.index("Thread Instructions Executed"); st=hdr.index("Warp Stall Sampling (All Samples)")
        d=data[kernel][(fileidx,int(r[0]))]
        d[0]+=float(r[ie] or 0); d[1]+=float(r[te] or 0); d[2]+=float(r[st] or 0); d[3]=r[1].strip()[:60]
want=sys.argv[1]
for k,dd in data.items():
    if want not in k: continue
    # identify the file block by its source text heuristics: print per-file totals
    files=collections.defaultdict(lambda:[0,0,0])
    for (f,l),v in dd.items():
        for i in range(3): files[f][i]+=v[i]
    tot=sum(v[0] for v in dd.values()); tst=sum(v[2] for v in dd.values())
    print(k[:60],'total inst',tot)
    for f,v in files.items():
        samp=[dd[(ff,l)][3] for (ff,l) in dd if ff==f][:2]
        print(' file',f,f"inst {100*v[0]/tot:.1f}% stall {100*v[2]/tst:.1f}% thr {v[1]/max(v[0],1):.1f}",samp)
    regions=[('coop_refine',53,135),('select_excl',180,214),('refine_mask',219,251),('refill',403,475),('prologue',476,533),('pool_core',573,603),('excl/memb task',604,628),('kind1 setup',628,681),('pool call',682,720),('select',720,756),('coop loop',756,782),('epilogue',782,880),('cta partial',140,173)]
    main=max(files,key=lambda f: sum(v[0] for (ff,l),v in dd.items() if ff==f and 403<=l<=880))
    for name,a,b in regions:
        s=[v for (f,l),v in dd.items() if f==main and a<=l<b]
        i=sum(v[0] for v in s); t=sum(v[1] for v in s); st=sum(v[2] for v in s)
        print(f'  {name:16s} inst {100*i/tot:5.1f}% stall {100*st/tst:5.1f}% thr {t/max(i,1):4.1f}')
print('--- device_util lines')
for k,dd in data.items():
    if want not in k: continue
    tot=sum(v[0] for v in dd.values()); tst=sum(v[2] for v in dd.values())
    for (f,l),v in sorted(dd.items(), key=lambda x:-x[1][0]):
        if f in (8,10) and v[0]/tot>0.003:
            print(f'  f{f} L{l:4d} inst {100*v[0]/tot:5.2f}% stall {100*v[2]/tst:5.2f}% thr {v[1]/max(v[0],1):4.1f} {v[3]}')
