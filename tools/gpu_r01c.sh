timeout 600 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
for q in K5-K2 K5-C4 K5-P5 K5-paw; do timeout 120 python tools/profile_query.py --part 0 --query $q --stats | cut -c1-220; done
for q in K1_4 C5 P5; do timeout 120 python tools/profile_query.py --part 1 --query $q --stats | cut -c1-220; done
