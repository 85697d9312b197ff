"""Aggregate ncu source-page warp-stall samples (tools/profile_stalls.sh) by CUDA source
line of K1<3,2,1>: python tools/stall_lines.py TAG CFG [N] (needs /tmp/sass/k1s3.sass from
nvdisasm -g of the same build)."""
import csv, gzip, re, sys
fn=None; line=None; off2line={}
for l in open('/tmp/sass/k1s3.sass'):
    m=re.match(r'\s*\.text\.(\S+):',l)
    if m: fn=m.group(1)
    m=re.search(r'//## File "([^"]+)", line (\d+)',l)
    if m: line=(m.group(1).split('/')[-1], int(m.group(2)))
    m=re.match(r'\s+/\*([0-9a-f]{4,})\*/',l)
    if m and fn and 'stream_kernelILi3ELi2ELi1E' in fn: off2line[int(m.group(1),16)]=line
tag=sys.argv[1]; cfg=sys.argv[2]; detail=len(sys.argv)>3
rows=list(csv.reader(gzip.open(f'gpurun_out/{tag}_{cfg}_source_sass.csv.gz','rt')))
hdr=rows[1]; data=rows[2:]
ia=hdr.index('Address'); iall=hdr.index('# Samples'); isrc=hdr.index('Source')
cols=[c for c in hdr if c.startswith('stall_') and '(Not' not in c]
base=int(data[0][ia],16)
agg={}
for r in data:
    try: off=int(r[ia],16)-base
    except: continue
    ln=off2line.get(off, ('?',0))
    key=ln if detail else ln[0]
    a=agg.setdefault(ln,{c:0 for c in cols+['all']})
    a['all']+=int(r[iall] or 0)
    for c in cols: a[c]+=int(r[hdr.index(c)] or 0)
src=open('/root/repo/paper_conf_ipps_leelv14_b200/csrc/arcv_device.cuh').read().split('\n')
tot=sum(a['all'] for a in agg.values()); print('total samples', tot)
for k,a in sorted(agg.items(), key=lambda x:-x[1]['all'])[:int(sys.argv[3]) if detail else 30]:
    top=sorted(((a[c],c) for c in cols), reverse=True)[:3]
    s=src[k[1]-1].strip()[:70] if k[0]=='arcv_device.cuh' else ''
    print(f"{a['all']:6d} {k[0][:22]:22s}:{k[1]:5d} {' '.join(f'{c[6:]}={v}' for v,c in top if v):50s} {s}")
