"""GPU parity of an index split past 2^31 (row f1; contraction.cpp split_large): an
outer product C[a,b] = A[a] B[b] with a = 3 * 2^30 BF16 elements (A 6.4 GB, C 19.3 GB) runs
as indices a (2^30 * 3/2) and a' (2).  Sampled a-values (random, the first and the last
ones, the split boundary) are compared bit-exactly with the CPU oracle on the gathered
sub-problem (the contraction is separable in a: each sampled row of C is the oracle's
"ab-a-b" over the gathered A values).  Needs a B200 with ~30 GB free: run with -m gpu."""
import numpy as np
import pytest
import torch

import oracle
import tcinputs
from paper_conf_cgo_kimstkpprs19_b200 import binding as tc
from paper_conf_cgo_kimstkpprs19_b200 import build

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module", autouse=True)
def _dev():
    if not torch.cuda.is_available():
        pytest.skip("no CUDA device")
    build.build()
    torch.cuda.set_device(0)


def test_outer_product_past_2_31():
    na, nb = 3 << 30, 3
    p = tc.plan("ab-a-b", f"a:{na};b:{nb}", dtype="bf16")
    names = {x["name"]: x["n"] for x in p.info()["indices"]}
    assert names == {"a": na // 2, "a'": 2, "b": nb}
    g = torch.Generator(device="cuda").manual_seed(7)
    A = torch.randint(-3, 4, (na,), generator=g, device="cuda", dtype=torch.int8).to(torch.bfloat16)
    B = torch.tensor([2.0, -3.0, 1.0], dtype=torch.bfloat16, device="cuda")
    C = torch.empty(na * nb, dtype=torch.bfloat16, device="cuda")
    p.execute(A, B, C)
    torch.cuda.synchronize()
    rng = np.random.default_rng(11)
    idx = np.unique(np.concatenate([rng.integers(0, na, 4096), np.arange(256), np.arange(na - 256, na),
                                    np.arange(na // 2 - 128, na // 2 + 128)]))
    ti = torch.from_numpy(idx).cuda()
    As = A[ti].cpu().view(torch.int16).numpy().view(np.uint16)
    Bs = B.cpu().view(torch.int16).numpy().view(np.uint16)
    got = C.view(nb, na)[:, ti].cpu().contiguous().view(torch.int16).numpy().view(np.uint16).reshape(-1)
    want = oracle.contract("ab-a-b", f"a:{idx.size};b:{nb}", As, Bs, dtype="bf16")
    bad = np.flatnonzero(got != want)
    assert bad.size == 0, (bad[:8], got[bad[:4]], want[bad[:4]])
    del A, C
    torch.cuda.empty_cache()
