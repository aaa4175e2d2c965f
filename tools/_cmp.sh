python tools/kprof.py lowrank 2>&1 | grep -v Warn | head -16
python tools/kprof.py factor 2>&1 | grep -v Warn | head -14
