import sys, re, csv, subprocess, collections
# usage: sassmap.py cubin fn_substr sass_csv srcfile
cubin, fsub, csvf, srcf = sys.argv[1:5]
dis = subprocess.run(['nvdisasm','-g','-c',cubin],capture_output=True,text=True).stdout.splitlines()
# find function section
infn=False; line=None; offs={}
for l in dis:
    if l.startswith('.text.') or re.match(r'\s*\.section\s+\.text\.',l):
        infn = fsub in l
        continue
    if not infn: continue
    m=re.search(r'//## File "(.*?)", line (\d+)',l)
    if m: line=(m.group(1).split('/')[-1],int(m.group(2))); continue
    m=re.match(r'\s*/\*([0-9a-f]{4,})\*/',l)
    if m and line is not None: offs[int(m.group(1),16)]=line
rows=list(csv.reader(open(csvf)))
h=rows[1]; data=rows[2:]
for i,r in enumerate(data):  # first kernel section only
    if r and r[0]=='Kernel Name': data=data[:i]; break
ia=h.index('Address'); ie=h.index('Instructions Executed'); iss=h.index('Warp Stall Sampling (All Samples)')
stalls=[i for i,n in enumerate(h) if n.startswith('stall_') and 'Not Issued' not in n]
base=int(data[0][ia],16)
agg=collections.defaultdict(lambda:[0,0,collections.Counter()])
tot_i=0; tot_s=0
for r in data:
    off=int(r[ia],16)-base
    ln=offs.get(off,-1)
    a=agg[ln]; ins=int(r[ie]); s=int(r[iss]); a[0]+=ins; a[1]+=s; tot_i+=ins; tot_s+=s
    for i in stalls:
        v=int(r[i]); 
        if v: a[2][h[i]]+=v
import os
srcs={}
def srcline(ln):
    if ln==-1: return ''
    f,n=ln
    if f not in srcs:
        p=os.path.join(os.path.dirname(srcf),f)
        srcs[f]=open(p).read().splitlines() if os.path.exists(p) else []
    L=srcs[f]
    return L[n-1].strip()[:70] if 0<n<=len(L) else ''
print('total inst',tot_i,'samples',tot_s, 'mapped offsets', len(offs))
for ln,(ins,s,c) in sorted(agg.items(), key=lambda kv:-kv[1][1])[:int(sys.argv[5]) if len(sys.argv)>5 else 40]:
    top=', '.join(f'{k[6:]}:{v}' for k,v in c.most_common(3))
    print(f'{str(ln):24s} inst {100*ins/tot_i:5.1f}% samp {100*s/tot_s:5.1f}%  [{top}]  {srcline(ln)}')
