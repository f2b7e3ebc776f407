import sys, time, faulthandler
faulthandler.enable()
sys.path.insert(0, ".")
import torch
torch.cuda.set_device(0)
import bench
print("pci", torch.cuda.get_device_properties(0).pci_bus_id, flush=True)
c = bench.ClockSampler(0)
c.start(); print("started", c.nvml is not None, flush=True)
x = torch.randn(4096, 4096, device="cuda")
for _ in range(200): x @ x
torch.cuda.synchronize(); time.sleep(0.5)
print(c.stop(), flush=True)
