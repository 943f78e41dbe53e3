"""Distinct CUDA streams for concurrency tests.

torch.cuda.Stream() hands out streams from a small recycled pool (32 per priority), so
"513 torch streams" are 32 CUDA streams.  These are real, separate cudaStream_t handles
(cuda-python runtime bindings), passed to the library as raw handles."""
from cuda.bindings import runtime as rt


class RawStream:
    def __init__(self):
        err, s = rt.cudaStreamCreateWithFlags(rt.cudaStreamNonBlocking)
        assert err == rt.cudaError_t.cudaSuccess, err
        self._s = s
        self.handle = int(s)

    def synchronize(self) -> None:
        err, = rt.cudaStreamSynchronize(self._s)
        assert err == rt.cudaError_t.cudaSuccess, err

    def query(self) -> bool:
        err, = rt.cudaStreamQuery(self._s)
        return err == rt.cudaError_t.cudaSuccess

    def destroy(self) -> None:
        if self._s is not None:
            rt.cudaStreamDestroy(self._s)
            self._s = None


def raw_streams(k: int) -> list:
    return [RawStream() for _ in range(k)]
