import sys, time
sys.path.insert(0, '.')
from paper_conf_ppopp_yehsser17_b200.pagoda import Pagoda, NO_START
from paper_conf_ppopp_yehsser17_b200 import tasks as T
with Pagoda(watchdog_s=5.0) as p:
    t0=time.time(); p.spawn_many(150000, 128, 1, 0, False, T.NOP, None); print("one session wrap ok", p.waitAll(), time.time()-t0, flush=True)
with Pagoda(watchdog_s=5.0, flags=NO_START) as p:
    for s in range(6):
        assert p.start() == 0
        try:
            p.spawn_many(30000, 128, 1, 0, False, T.NOP, None)
        except Exception as e:
            print("session", s, "spawn failed", e, p.counters(), flush=True); break
        print("session", s, "stop", p.stop(), flush=True)
with Pagoda(watchdog_s=5.0, flags=NO_START) as p:
    for s in range(6):
        assert p.start() == 0
        try:
            p.spawn_many(30000, 128, 1, 2048, True, T.NOP, None)
        except Exception as e:
            print("shmem session", s, "spawn failed", e, flush=True); break
        print("shmem session", s, "stop", p.stop(), flush=True)
