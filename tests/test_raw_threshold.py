"""The fused kernels test the headroom on the output accumulator before its
fp32 bias (y_raw <= T with T = raw_threshold(H, b4)); this host test checks
that the test decides exactly what fl(y_raw + b4) <= H decides
(tests/cpp/raw_threshold_test.cu, compiled with nvcc against the library's
own device_common.cuh; no GPU)."""
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def test_raw_threshold_equivalence(tmp_path):
    src = os.path.join(ROOT, "tests", "cpp", "raw_threshold_test.cu")
    exe = str(tmp_path / "raw_threshold_test")
    subprocess.check_call([NVCC, "-std=c++17", "-O1", "-gencode", "arch=compute_100a,code=sm_100a", "-o", exe, src])
    out = subprocess.run([exe], capture_output=True, text=True)
    assert out.returncode == 0, out.stdout + out.stderr
    assert "ok" in out.stdout
