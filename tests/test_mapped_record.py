"""Host-side protocol of the host-mapped decision record (no GPU): a complete
record is accepted for its own sequence number only; stale, partially
written, torn and corrupted records are refused (tests/cpp/mapped_record_test.cu
compiled with nvcc against the library's own common.cuh)."""
import os
import subprocess

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
NVCC = os.environ.get("NVCC", "/usr/local/cuda/bin/nvcc")


def test_mapped_record_protocol(tmp_path):
    src = os.path.join(ROOT, "tests", "cpp", "mapped_record_test.cu")
    exe = str(tmp_path / "mapped_record_test")
    subprocess.check_call([NVCC, "-std=c++17", "-O1", "-o", exe, src])
    out = subprocess.run([exe], capture_output=True, text=True)
    assert out.returncode == 0, out.stderr
    assert "ok" in out.stdout
