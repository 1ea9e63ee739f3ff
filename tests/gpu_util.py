"""Helpers for the GPU parity tests: put a host word array on the device at a
chosen misalignment, surrounded by canary words, and bring the WHOLE buffer
(canaries included) back for a bit-exact comparison with the oracle."""
import numpy as np
import torch

PRE = 16          # canary words before the buffer (plus the misalignment)
POST = 16         # canary words after the buffer's capacity
CANARY = 0xC0FFEE00


def canaries(k):
    return (np.arange(k, dtype=np.uint32) + CANARY).astype(np.uint32)


class DevBuf:
    """Device copy of `host` (uint32 words) starting `mis` words past a
    16-byte boundary, with `capacity >= host.size` words of room."""

    def __init__(self, host, mis=0, capacity=None, device="cuda"):
        host = np.ascontiguousarray(host, dtype=np.uint32)
        self.n = host.size
        self.cap = capacity if capacity is not None else self.n
        self.pre = PRE + mis
        total = self.pre + self.cap + POST
        full = np.empty(total, dtype=np.uint32)
        full[:self.pre] = canaries(self.pre)
        full[self.pre:self.pre + self.n] = host
        full[self.pre + self.n:self.pre + self.cap] = 0x5EED5EED
        full[self.pre + self.cap:] = canaries(POST) + 0x100
        self.expected_full = full.copy()
        self.t = torch.from_numpy(full.view(np.int32)).to(device)
        assert self.t.data_ptr() % 16 == 0

    @property
    def ptr(self):
        return self.t.data_ptr() + 4 * self.pre

    def host_region(self):
        """Copy of the initial content of [ptr, ptr + cap)."""
        return self.expected_full[self.pre:self.pre + self.cap].copy()

    def fetch(self):
        torch.cuda.synchronize()
        return self.t.cpu().numpy().view(np.uint32)

    def assert_equals(self, expected_region, what=""):
        got = self.fetch()
        exp = self.expected_full.copy()
        exp[self.pre:self.pre + self.cap] = expected_region
        if not np.array_equal(got, exp):
            bad = np.nonzero(got != exp)[0]
            i = int(bad[0])
            raise AssertionError(
                f"{what}: {bad.size} words differ; first at buffer word {i - self.pre} "
                f"(got {got[i]:#x}, expected {exp[i]:#x}); canary region: "
                f"{'yes' if i < self.pre or i >= self.pre + self.cap else 'no'}")
