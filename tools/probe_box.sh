nproc; free -g; lscpu | head -20; nvidia-smi; nvidia-smi topo -m; nvidia-smi -q | grep -i -A3 "pcie\|link width\|Max" | head -60
python - <<'PY'
import torch,time
d=torch.device('cuda:0')
print(torch.cuda.get_device_properties(0))
for sz in [1<<20, 16<<20, 256<<20, 1<<30]:
    h=torch.empty(sz,dtype=torch.uint8).pin_memory(); g=torch.empty(sz,dtype=torch.uint8,device=d)
    s=torch.cuda.Stream()
    best=0
    for i in range(5):
        e0=torch.cuda.Event(enable_timing=True); e1=torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            e0.record(); g.copy_(h,non_blocking=True); e1.record()
        e1.synchronize(); t=e0.elapsed_time(e1)/1e3; best=max(best,sz/t/1e9)
    print("H2D",sz,best,"GB/s")
    best=0
    for i in range(5):
        e0=torch.cuda.Event(enable_timing=True); e1=torch.cuda.Event(enable_timing=True)
        with torch.cuda.stream(s):
            e0.record(); h.copy_(g,non_blocking=True); e1.record()
        e1.synchronize(); t=e0.elapsed_time(e1)/1e3; best=max(best,sz/t/1e9)
    print("D2H",sz,best,"GB/s")
PY
