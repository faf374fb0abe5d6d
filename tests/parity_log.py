"""Achieved-error recorder of the GPU parity tests (VERDICT r1 "parity hardening").

Every `_check` in tests/test_gpu_parity.py reports, per output tensor, the normwise
max|gpu − ref| / max|ref| (the judged bf16 metric, reading R19), the RMS-relative error
‖gpu − ref‖₂ / ‖ref‖₂ and the max abs error.  At session end tests/conftest.py writes them to
gpurun_out/parity_errors.jsonl (one JSON object per tensor); DESIGN.md §3 summarises them."""
RECORDS = []


def record(ctx, key, dtype, normwise, rms_rel, max_abs, tol):
    RECORDS.append({"ctx": ctx, "tensor": key, "dtype": dtype, "normwise_rel": normwise,
                    "rms_rel": rms_rel, "max_abs": max_abs, "tol": tol})
