timeout 900 python tools/qos_tail.py --queries 10000 --policy baymax 2>&1 | tail -8
