"""Probe cudaHostRegister of /dev/shm mappings of growing size (multi-process host table)."""
import mmap, os, time, sys
import numpy as np, torch
torch.cuda.init()
cr = torch.cuda.cudart()
for gb in [int(x) for x in sys.argv[1:]]:
    n = gb << 30
    path = f"/dev/shm/gd_probe_{gb}"
    with open(path, "wb") as f:
        f.truncate(n)
    fd = os.open(path, os.O_RDWR)
    mm = mmap.mmap(fd, n, mmap.MAP_SHARED, mmap.PROT_READ | mmap.PROT_WRITE)
    os.close(fd)
    a = np.frombuffer(mm, dtype=np.uint8)
    t = torch.from_numpy(a)
    t0 = time.time()
    touch = os.environ.get("TOUCH") == "1"
    if touch:
        t.view(-1)[::4096].fill_(1)
    t1 = time.time()
    rc = cr.cudaHostRegister(t.data_ptr(), n, 3)
    t2 = time.time()
    print(f"{gb} GB: touch={touch} {t1-t0:.1f}s register rc={int(rc)} {t2-t1:.1f}s", flush=True)
    if int(rc) == 0:
        cr.cudaHostUnregister(t.data_ptr())
    del t, a
    mm.close()
    os.unlink(path)
