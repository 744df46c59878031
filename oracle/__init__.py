"""CPU float64 oracle — TEST INFRASTRUCTURE ONLY (see fmmfft_oracle.py's header).
Only tests/, __graft_entry__.smoke() and bench.py's cpu_baseline / --impl reference legs import it."""
