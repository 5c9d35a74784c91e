import sys, time, os
sys.path.insert(0, os.getcwd())
import torch
from paper_conf_icppw_tiancd23_b200 import Args, workloads, _ens
name = sys.argv[1]
if name == "C2U":
    lines = [l.replace("-G hash -h 10000", "-G unionized") for l in workloads.c2(24)]
else:
    lines = workloads.tstar(1024)
args = Args.parse(workloads.text(lines))
cfg = _ens.make_cfg(len(lines), threads=512)
t = time.perf_counter(); ws = _ens.workspace_bytes("auto", args, cfg); print("workspace_bytes %.1f ms" % ((time.perf_counter() - t) * 1e3), ws / 1e9, "GB")
buf = torch.empty(ws, dtype=torch.uint8, device="cuda")
stream = torch.cuda.current_stream().cuda_stream
for it in range(3):
    torch.cuda.synchronize()
    t0 = time.perf_counter(); run = _ens.Run.launch("auto", args, cfg, buf.data_ptr(), ws, stream, keep=buf)
    t1 = time.perf_counter(); torch.cuda.synchronize()
    t2 = time.perf_counter(); out = run.collect()
    t3 = time.perf_counter(); run.close()
    t4 = time.perf_counter()
    print("launch %.1f  kernel-wait %.1f  collect %.1f  close %.1f ms" % ((t1-t0)*1e3, (t2-t1)*1e3, (t3-t2)*1e3, (t4-t3)*1e3), flush=True)
