"""TEST INFRASTRUCTURE ONLY: the CPU oracle (see oracle.h).  Only tests/, smoke() and
bench.py's cpu_baseline / --impl reference leg may import it."""
