#!/bin/bash
bash tools/gpurun/run62.sh
bash tools/gpurun/run63.sh
