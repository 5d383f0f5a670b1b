import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_sunlyjlq22_b200 as sm, stencil_inputs as si
acc, c = si.heat3d()
p = sm.Plan((64, 64, 64), acc, c, "f64", "ST_RT_PR")
uid = sm.nccl_unique_id()
try:
    p.set_comm(uid, 0, 1)
    print("set_comm ok, ghost", p.ghost)
except Exception as e:
    print("ERR", e)
import torch.distributed as dist
os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT="29555", RANK="0", WORLD_SIZE="1")
dist.init_process_group("nccl", device_id=torch.device("cuda", 0))
t = torch.ones(4, device="cuda"); dist.all_reduce(t); torch.cuda.synchronize()
be = dist.distributed_c10d._get_default_group()._get_backend(torch.device("cuda"))
print("torch nccl ok", t.tolist(), hasattr(be, "_comm_ptr"))
try:
    print("comm ptr", be._comm_ptr())
except Exception as e:
    print("comm_ptr ERR", e)
