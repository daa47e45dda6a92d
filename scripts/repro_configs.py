import os, sys, json
sys.path.insert(0, os.getcwd())
import torch
import bench
import paper_conf_ipps_awasthillw16_b200 as lib
dev = torch.device("cuda", 0)
stream = torch.cuda.current_stream(dev)
out = bench.bench_configs(lib, dev, stream)
print(json.dumps(out)[:3000])
