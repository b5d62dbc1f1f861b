"""The device input generator (libsynth) is bit-identical to the numpy generator."""
import numpy as np
import pytest

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu
if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import synth
import synth.gpu as SG

DEV = torch.device("cuda", 0)


@pytest.mark.parametrize("mode,wdtype,dim", [("float", "f32", 64), ("float", "bf16", 256), ("int", "f32", 16),
                                             ("identity", "f32", 8), ("identity", "bf16", 32)])
def test_tables_bitexact(mode, wdtype, dim):
    w = synth.make_workload("tiny", G=1, mode=mode, wdtype=wdtype, odtype=wdtype, dim=dim, rows=5000)
    Wd = SG.gen_table(w, 3, 5000, DEV)
    torch.cuda.synchronize()
    ref = synth.table_rows(w.table_seed, 3, 5000, dim, mode, wdtype)
    if wdtype == "bf16":
        got = Wd.view(torch.int16).cpu().numpy().view(np.uint16)
        assert np.array_equal(got, synth.to_bf16_bits(ref))
    else:
        assert np.array_equal(Wd.cpu().numpy().view(np.uint32), ref.view(np.uint32))


@pytest.mark.parametrize("name,G,r,over", [("tiny", 2, 1, dict(pmin=0, pmax=40, B=999, dist="zipf", rows=12345)),
                                           ("tiny", 1, 0, dict(pmin=1, pmax=128, B=3000, T=3, dist="uniform")),
                                           ("single", 1, 0, dict(T=2))])
def test_csr_bitexact(name, G, r, over):
    w = synth.make_workload(name, G=G, **over)
    o_d, x_d = SG.rank_csr(w, 4242, r, DEV)
    o, x = synth.rank_csr(w, 4242, r)
    assert np.array_equal(o_d.cpu().numpy(), o)
    assert np.array_equal(x_d.cpu().numpy(), x)


def test_large_table_rows_sampled():
    w = synth.make_workload("weak", G=1)
    W = SG.gen_table(w, 7, 2_000_000, DEV)
    rows = np.array([0, 1, 999_999, 1_999_999, 123_457])
    got = W[torch.from_numpy(rows).to(DEV)].cpu().numpy()
    assert np.array_equal(got.view(np.uint32), synth.table_values(w.table_seed, 7, rows, 128).view(np.uint32))
