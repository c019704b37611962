#!/bin/bash
./tools/gpu_round.sh "$@"
./tools/gpu_profile.sh
