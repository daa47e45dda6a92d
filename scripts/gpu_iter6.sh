mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_sa.py tests/test_gpu_sync.py tests/test_gpu_sa_init.py -x -q > gpurun_out/pytest_iter.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/pytest_iter.log
cat > /tmp/t500.py <<'PY'
import os, sys, torch
sys.path.insert(0, os.getcwd())
import gen, paper_conf_ipps_awasthillw16_b200 as cdd
for n in (300, 500):
    ins = cdd.Instance.from_gen(gen.cdd_instance(n, 1, 0.6))
    C, S = 65536, 1000
    for env in ("0", "1"):
        if env == "1": os.environ["CDD_SA_NO_NIB"] = "1"
        ws = cdd.sa_run(ins, C, S, seed=1, T0=1000.0)["workspace"]
        torch.cuda.synchronize()
        e1, e2 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e1.record(); cdd.sa_run(ins, C, S, seed=1, T0=1000.0, workspace=ws); e2.record(); torch.cuda.synchronize()
        print(n, "byte rows" if env == "1" else "small-weight", cdd.sa_layout(ins, C), C * (S + 1) / (e1.elapsed_time(e2) / 1000))
        os.environ.pop("CDD_SA_NO_NIB", None)
PY
python /tmp/t500.py
