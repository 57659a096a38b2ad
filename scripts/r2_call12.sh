#!/bin/bash
bash scripts/r2_call10.sh
bash scripts/r2_call11.sh
