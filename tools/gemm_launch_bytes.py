# per-GEMM DRAM bytes / time of one FLUX 2048^2 step from an ncu launch list: python tools/gemm_launch_bytes.py <launches.csv>
import csv,sys,collections
def load(f):
    rows=list(csv.reader(open(f)))
    hi=[i for i,r in enumerate(rows) if "Kernel Name" in r][0]; h=rows[hi]
    ii,ki,mi,vi,ui=(h.index(c) for c in ("ID","Kernel Name","Metric Name","Metric Value","Metric Unit"))
    sc={"byte":1,"Kbyte":1e3,"Mbyte":1e6,"Gbyte":1e9,"nsecond":1,"usecond":1e3,"msecond":1e6}
    per=collections.OrderedDict()
    for r in rows[hi+1:]:
        if len(r)<=vi: continue
        d=per.setdefault(r[ii],{"name":r[ki][:40]})
        d[r[mi]]=float(r[vi].replace(",",""))*sc.get(r[ui],1)
    return list(per.values())
L=load(sys.argv[1])
g=[d for d in L if "gemm" in d["name"]]
# double blocks: 19 x 4 gemms, singles: 38 x 2
names=["qkv","proj","fc1","fc2"]*19+["lin1","lin2"]*38
agg=collections.defaultdict(lambda:[0,0,0])
for d,n in zip(g[1:],names):   # first gemm = img_in? check count
    a=agg[n]; a[0]+=1; a[1]+=d["dram__bytes_read.sum"]+d["dram__bytes_write.sum"]; a[2]+=d["gpu__time_duration.sum"]
print(len(g))
for n,(c,b,t) in agg.items(): print(n, c, round(b/c/1e6,1),"MB", round(t/c/1e3,1),"us")
