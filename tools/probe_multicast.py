"""Probe: NVSwitch multicast support and torch symmetric-memory rendezvous on
this box (world size from the environment, default 1)."""
import os
import torch
import torch.distributed as dist
import torch.distributed._symmetric_memory as symm_mem
from cuda.bindings import driver as drv

os.environ.setdefault("MASTER_ADDR", "127.0.0.1")
os.environ.setdefault("MASTER_PORT", "29533")
os.environ.setdefault("RANK", "0")
os.environ.setdefault("WORLD_SIZE", "1")
torch.cuda.set_device(int(os.environ.get("LOCAL_RANK", "0")))
drv.cuInit(0)
err, dev = drv.cuDeviceGet(torch.cuda.current_device())
err, mc = drv.cuDeviceGetAttribute(drv.CUdevice_attribute.CU_DEVICE_ATTRIBUTE_MULTICAST_SUPPORTED, dev)
print("multicast supported attr:", err, mc, flush=True)
dist.init_process_group("nccl", device_id=torch.device("cuda", torch.cuda.current_device()))
try:
    t = symm_mem.empty(64, dtype=torch.int64, device="cuda")
    h = symm_mem.rendezvous(t, dist.group.WORLD.group_name)
    print("rendezvous ok; multicast_ptr", hex(h.multicast_ptr), "buffer_ptrs", [hex(p) for p in h.buffer_ptrs],
          "signal", [hex(p) for p in h.signal_pad_ptrs][:2], flush=True)
    t.fill_(3)
    h.barrier()
    torch.cuda.synchronize()
    print("barrier ok", flush=True)
except Exception as e:  # noqa: BLE001
    print("symm_mem failed:", repr(e)[:400], flush=True)
dist.destroy_process_group()
