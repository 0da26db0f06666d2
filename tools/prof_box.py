import sys, torch
sys.path.insert(0, ".")
import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_torch
r = int(sys.argv[1]) if len(sys.argv) > 1 else 4
u8 = make_torch(1080, 1920, "int32", "u8", seed=5, batch=32, device="cuda").to(torch.uint8)
box = torch.empty(32, 1080, 1920, dtype=torch.int32, device="cuda")
for _ in range(3):
    libsat.box_filter(u8, r, r, out=box)
torch.cuda.synchronize()
