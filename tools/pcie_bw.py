import torch, time
d=torch.device('cuda',0)
for mb in [1,8,17,64]:
    n=mb<<20
    h=torch.empty(n,dtype=torch.uint8).pin_memory(); g=torch.empty(n,dtype=torch.uint8,device=d)
    for _ in range(3): g.copy_(h,non_blocking=True); h.copy_(g,non_blocking=True)
    torch.cuda.synchronize()
    s=torch.cuda.Event(enable_timing=True); e=torch.cuda.Event(enable_timing=True)
    s.record(); 
    for _ in range(10): g.copy_(h,non_blocking=True)
    e.record(); torch.cuda.synchronize(); t1=s.elapsed_time(e)/10
    s.record()
    for _ in range(10): h.copy_(g,non_blocking=True)
    e.record(); torch.cuda.synchronize(); t2=s.elapsed_time(e)/10
    # concurrent both directions on two streams
    s1=torch.cuda.Stream(); s2=torch.cuda.Stream(); h2=torch.empty(n,dtype=torch.uint8).pin_memory(); g2=torch.empty(n,dtype=torch.uint8,device=d)
    torch.cuda.synchronize(); t0=time.perf_counter()
    for _ in range(10):
        with torch.cuda.stream(s1): g.copy_(h,non_blocking=True)
        with torch.cuda.stream(s2): h2.copy_(g2,non_blocking=True)
    torch.cuda.synchronize(); t3=(time.perf_counter()-t0)/10*1e3
    print(f"{mb} MB: H2D {mb/1024/t1*1e3:.1f} GB/s  D2H {mb/1024/t2*1e3:.1f} GB/s  both-dir per pair {t3:.3f} ms ({2*mb/1024/t3*1e3:.1f} GB/s agg)")
