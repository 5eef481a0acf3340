# L56 timing of experiment builds (BQR lib override) + parity of the LU tests
for lib in "$@"; do
python - "$lib" <<'PY'
import sys, os, json
sys.path.insert(0, os.getcwd())
import paper_conf_ipps_andersonsk12_b200 as bqr
bqr._LIB_PATH = os.path.abspath(sys.argv[1])
import torch, bench
w = bench.Workload("L56", 0, 1, torch, bqr)
flush = torch.empty(256 << 20, dtype=torch.uint8, device="cuda")
_, q = bench.time_workload(w, 50, 5, torch, None, 1, flush)
print(json.dumps({"lib": sys.argv[1], "L56_us": round(q * 1e3, 2)}))
PY
done
