import sys, os, json, torch
sys.path.insert(0, '/root/repo')
import bench
import paper_conf_pldi_dubachcrbf12_b200 as lime
lime.load()
flush = torch.empty(2 * torch.cuda.get_device_properties(0).L2_cache_size, dtype=torch.uint8, device="cuda")
x = torch.ones(1 << 20, device="cuda"); out = torch.empty(1, device="cuda")
f = lambda: lime.reduce_sum(x[:1], out=out)
def plain(fn, it=50):
    for _ in range(5): fn()
    torch.cuda.synchronize(); r=[]
    for _ in range(it):
        a,b=torch.cuda.Event(enable_timing=True),torch.cuda.Event(enable_timing=True)
        a.record(); fn(); b.record(); torch.cuda.synchronize(); r.append(a.elapsed_time(b)*1e3)
    r.sort(); return r[len(r)//2]
def sleep_only(fn, it=50):
    for _ in range(5): fn()
    torch.cuda.synchronize(); ev=[]
    for _ in range(it):
        a,b=torch.cuda.Event(enable_timing=True),torch.cuda.Event(enable_timing=True)
        torch.cuda._sleep(bench.SLEEP_CYCLES); a.record(); fn(); b.record(); ev.append((a,b))
    torch.cuda.synchronize(); r=sorted(a.elapsed_time(b)*1e3 for a,b in ev); return r[len(r)//2]
def empty_pair(it=50):
    r=[]
    for _ in range(it):
        a,b=torch.cuda.Event(enable_timing=True),torch.cuda.Event(enable_timing=True)
        torch.cuda._sleep(bench.SLEEP_CYCLES); a.record(); b.record(); torch.cuda.synchronize(); r.append(a.elapsed_time(b)*1e3)
    r.sort(); return r[len(r)//2]
def graph_per_launch(fn, k=200):
    g=torch.cuda.CUDAGraph(); s=torch.cuda.Stream()
    with torch.cuda.stream(s):
        fn(); torch.cuda.synchronize()
        with torch.cuda.graph(g):
            for _ in range(k): fn()
    g.replay(); torch.cuda.synchronize()
    a,b=torch.cuda.Event(enable_timing=True),torch.cuda.Event(enable_timing=True)
    a.record(); g.replay(); b.record(); torch.cuda.synchronize(); return a.elapsed_time(b)*1e3/k
res={"event_pair_only_us": empty_pair(),
     "reduce_1elem_plain_us": plain(f), "reduce_1elem_sleep_us": sleep_only(f),
     "reduce_1elem_flush_sleep_us": bench.time_launches(f, 50, 5, flush)[0]*1e3,
     "reduce_1elem_graph_per_launch_us": graph_per_launch(f)}
print(json.dumps(res))
