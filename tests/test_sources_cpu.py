"""Source hygiene: no file that travels to the GPU box names a copy call the GPU pool has
closed (the batched memcpy family raised Xid 32 faults there; gpurun refuses a snapshot
whose sources name it).  Notes (.md) may mention it."""
import os

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
CLOSED = ["Memcpy" + "BatchAsync", "Memcpy3D" + "BatchAsync"]
SKIP_DIRS = {".git", "gpurun_out", "__pycache__", ".pytest_cache", "baseline", "profiles"}
SOURCE_EXT = (".cu", ".cuh", ".cc", ".cpp", ".c", ".h", ".py", ".sh")


def test_no_closed_copy_calls_in_sources():
    hits = []
    for dirpath, dirnames, filenames in os.walk(ROOT):
        dirnames[:] = [d for d in dirnames if d not in SKIP_DIRS]
        for f in filenames:
            if not f.endswith(SOURCE_EXT):
                continue
            path = os.path.join(dirpath, f)
            with open(path, errors="replace") as fh:
                text = fh.read()
            hits += [f"{os.path.relpath(path, ROOT)}: {name}" for name in CLOSED if name in text]
    assert not hits, hits
