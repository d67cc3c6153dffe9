#!/bin/bash
timeout 600 python scripts/ab_xs.py
LARGE=1 timeout 600 python scripts/ab_xs.py
