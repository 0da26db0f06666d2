import sys, torch
sys.path.insert(0, ".")
import paper_conf_icpp_kasagini14_b200 as libsat
from sat_inputs import make_torch
v = sys.argv[1]
x = make_torch(16384, 16384, "int32", "u32", seed=1, device="cuda")
y = torch.empty_like(x)
for _ in range(3):
    libsat.sat(x, variant=v, out=y)
torch.cuda.synchronize()
print("launches", libsat.last_launch_count(), "r_eff", libsat.last_r_effective())
