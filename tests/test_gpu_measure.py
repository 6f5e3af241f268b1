"""The measurement helpers bench.py builds its roofline on (include/dycuckoo.h,
"Measurement helpers"): the random-bucket gather and its read-then-store
variant.  They are not part of the method; these checks only make sure the
ceilings they report come from kernels that really touch the buffer."""
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

from paper_conf_icde_lizlhs21_b200 import _lib as L  # noqa: E402


@pytest.mark.parametrize("bytes_per_read", [32, 64, 128, 256])
def test_gather_reads_leave_buffer_and_writes_change_it(bytes_per_read):
    buf = torch.zeros(1 << 22, dtype=torch.uint8, device="cuda")
    sink = torch.zeros(1, dtype=torch.int64, device="cuda")
    s = torch.cuda.current_stream().cuda_stream
    L.check(L.dyc_bench_gather(buf.data_ptr(), buf.numel(), 1 << 16, bytes_per_read, 7, sink.data_ptr(), s), "gather")
    torch.cuda.synchronize()
    assert int(buf.count_nonzero()) == 0, "the read-only gather must not write"
    L.check(L.dyc_bench_gather_ex(buf.data_ptr(), buf.numel(), 1 << 16, bytes_per_read, 7, L.DYC_GATHER_WRITE,
                                  sink.data_ptr(), s), "gather_ex")
    torch.cuda.synchronize()
    words = buf.view(torch.int64)
    touched = int((words != 0).sum())
    units = buf.numel() // bytes_per_read
    # one 8-byte store per read into the bucket read: at most 2^16 words, and
    # (2^16 reads over `units` buckets) most of the distinct buckets drawn
    assert 0 < touched <= 1 << 16
    assert touched >= min(units, 1 << 16) // 4


def test_gather_rejects_bad_arguments():
    buf = torch.zeros(1 << 16, dtype=torch.uint8, device="cuda")
    sink = torch.zeros(1, dtype=torch.int64, device="cuda")
    s = torch.cuda.current_stream().cuda_stream
    assert L.dyc_bench_gather(buf.data_ptr(), buf.numel(), 16, 48, 1, sink.data_ptr(), s) == L.DYC_ERR_INVALID_ARG
    assert L.dyc_bench_gather_ex(buf.data_ptr(), buf.numel(), 16, 64, 1, 8, sink.data_ptr(), s) == L.DYC_ERR_INVALID_ARG
    assert L.dyc_bench_gather(buf.data_ptr(), 16, 16, 64, 1, sink.data_ptr(), s) == L.DYC_ERR_INVALID_ARG
