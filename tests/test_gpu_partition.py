"""SM partition (green contexts, wind_kv_partition_sms): disjoint SM
sets for the migration and for co-running compute.  An op on the migration stream is
byte-exact vs the oracle and completes; torch work runs on the compute stream; the SM
counts add up to the device's."""
import numpy as np
import pytest
import torch

import oracle as O
import paper_conf_isca_fenghzly025_b200 as wk

pytestmark = pytest.mark.gpu


def test_partition_streams_run_a_migration_and_compute():
    sms = torch.cuda.get_device_properties(0).multi_processor_count
    P = wk.Partition(0, 8)
    try:
        assert P.sms_migration >= 8 and P.sms_migration % 8 == 0
        assert P.sms_migration + P.sms_compute <= sms and P.sms_compute > 0
        L, H, d, bs, eb = 4, 8, 128, 16, 2
        src = wk.Pool(L, H, d, bs, eb, 300)
        dst = wk.Pool(L, H, d, bs, eb, 320)
        rng = np.random.default_rng(0)
        s0 = rng.integers(0, 256, src.nbytes, dtype=np.uint8)
        d0 = rng.integers(0, 256, dst.nbytes, dtype=np.uint8)
        src.tensor().copy_(torch.from_numpy(s0))
        dst.tensor().copy_(torch.from_numpy(d0))
        torch.cuda.synchronize()
        sbt = rng.permutation(300)[:250].astype(np.int32)
        dbt = rng.permutation(320)[:250].astype(np.int32)
        ts, td = torch.as_tensor(sbt, device="cuda"), torch.as_tensor(dbt, device="cuda")
        torch.cuda.synchronize()
        wk.migrate(src, ts, dst, td, stream=P.migration)
        t = dst.layer_ticket()
        wk.layer_wait(dst, L - 1, t, stream=P.compute)      # compute partition waits on the flag
        with torch.cuda.stream(P.compute):
            x = torch.ones(1 << 20, device="cuda") * 3.0
            y = (x * 2).sum()
        torch.cuda.synchronize()
        assert float(y) == 6.0 * (1 << 20)
        want = d0.copy()
        g = lambda p: O.Geom(0, L, H, d, bs, eb, p.desc.n_blocks)  # noqa: E731
        assert O.migrate(s0, g(src), sbt, want, g(dst), dbt, 0, L) == O.OK
        np.testing.assert_array_equal(dst.tensor().cpu().numpy(), want)
    finally:
        torch.cuda.synchronize()
        P.destroy()


def test_partition_rejects_bad_arguments():
    with pytest.raises(wk.WindKVError):
        wk.Partition(0, 0)
    with pytest.raises(wk.WindKVError):
        wk.Partition(0, 100000)
