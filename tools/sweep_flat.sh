for cfg in "4 16" "1 16" "1 64" "1 256" "2 64" "1 1024"; do set -- $cfg
  echo "units/cta=$1 min_rounds=$2"
  XR_FLAT_UNITS_PER_CTA=$1 XR_FLAT_MIN_ROUNDS=$2 python - <<'PY'
import sys, os, json, torch
sys.path.insert(0, os.getcwd())
import paper_conf_ppopp_xutycc14_b200 as xr
for dims, lv, dt, tdt in [((1 << 20, 2, 32), "g", "int32", torch.int32), ((1 << 20, 2, 32), "g", "fp64", torch.float64),
                          ((512, 512, 512), "gw", "int32", torch.int32)]:
    n = dims[0] * dims[1] * dims[2]
    x = torch.ones(n, dtype=tdt, device="cuda"); o = torch.zeros(xr.xr_out_count(dims, lv), dtype=tdt, device="cuda")
    for _ in range(3): xr.xr_reduce("+", dt, dims, lv, x.data_ptr(), o.data_ptr())
    torch.cuda.synchronize(); a, b = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    a.record()
    for _ in range(10): xr.xr_reduce("+", dt, dims, lv, x.data_ptr(), o.data_ptr())
    b.record(); torch.cuda.synchronize(); ms = a.elapsed_time(b) / 10
    p = xr.xr_plan_describe("+", dt, dims, lv, x.data_ptr())
    print("  ", dims, lv, dt, p["kernel"], p["units"], round(ms * 1e3, 1), "us", round(n * x.element_size() / ms / 1e6), "GB/s")
PY
done
