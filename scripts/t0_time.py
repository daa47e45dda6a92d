import sys; sys.path.insert(0,'.')
import torch, gen, paper_conf_ipps_awasthillw16_b200 as cdd
ins = cdd.Instance.from_gen(gen.cdd_instance(1000, 1, 0.4))
for _ in range(3): cdd.sa_t0(ins, samples=5000)
torch.cuda.synchronize()
