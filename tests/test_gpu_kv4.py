"""GPU parity of NEXT-4 (INT4 KV cache; reading R17) through the C ABI:
codes, scales and mins bit-exact against the oracle; the dequantised tensor bit-exact against
the oracle's binary32 dequantisation rounded to f16/bf16."""
import numpy as np
import pytest

from oracle import kv4 as okv
from paper_conf_asplos_liu0rxpwl0w25_b200 import synth

torch = pytest.importorskip("torch")
pytestmark = pytest.mark.gpu

if not torch.cuda.is_available():
    pytest.skip("no CUDA device", allow_module_level=True)

import paper_conf_asplos_liu0rxpwl0w25_b200 as cb   # noqa: E402

DEV = "cuda:0"


@pytest.mark.parametrize("T,C,G,bf16", [
    (1, 64, 32, False), (37, 128, 32, False), (300, 1024, 128, True), (4096, 1024, 128, False),
    (513, 512, 256, False), (100, 192, 64, True),
])
def test_kv4_parity(T, C, G, bf16):
    rng = np.random.default_rng(T + C + G)
    x = synth.make_kv(T, C, rng, bf16=bf16)
    xf = synth.bf16_bits_to_f32(x) if bf16 else x.astype(np.float32)
    xd = torch.from_numpy(x.view(np.int16)).to(DEV).view(torch.bfloat16) if bf16 else torch.from_numpy(x).to(DEV)
    codes, scales, mins = cb.kv4_quantize(xd, G)
    out_dt = torch.bfloat16 if bf16 else torch.float16
    y = cb.kv4_dequantize(codes, scales, mins, G, out_dtype=out_dt)
    torch.cuda.synchronize()
    q, s, mn = okv.quantize(xf, G)
    assert np.array_equal(codes.cpu().numpy(), okv.pack(q)), "codes differ"
    assert np.array_equal(scales.cpu().numpy().view(np.uint32), s.view(np.uint32)), "scales differ"
    assert np.array_equal(mins.cpu().numpy().view(np.uint32), mn.view(np.uint32)), "mins differ"
    ref = okv.dequantize(q, s, mn, G)
    ref_t = torch.from_numpy(ref).to(out_dt)
    assert torch.equal(y.cpu().view(torch.int16), ref_t.view(torch.int16)), "dequantised values differ"


def test_kv4_strided_input():
    rng = np.random.default_rng(5)
    x = synth.make_kv(200, 256, rng)
    big = torch.zeros((200, 320), dtype=torch.float16, device=DEV)
    big[:, :256] = torch.from_numpy(x).to(DEV)
    codes, scales, mins = cb.kv4_quantize(big[:, :256], 64)
    torch.cuda.synchronize()
    q, s, mn = okv.quantize(x.astype(np.float32), 64)
    assert np.array_equal(codes.cpu().numpy(), okv.pack(q))
