"""CPU oracle for the A-ABFT hot path -- TEST INFRASTRUCTURE ONLY (see oracle.py header)."""
